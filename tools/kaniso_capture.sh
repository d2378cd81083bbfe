cd /root/repo
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
MAS_NO_GRAPH=1 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_aniso --launch-skip 3 --launch-count 1 -f -o gpurun_out/r3c_C2a_kaniso python tools/prof_driver.py --config C2a > gpurun_out/r3c_kaniso.log 2>&1
echo rc=$?
