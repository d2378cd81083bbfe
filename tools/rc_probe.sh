#!/bin/bash
# racecheck / synccheck probes of the graph-loop residue (round 2)
cd "$(dirname "$0")/.."
O=gpurun_out; CS=/usr/local/cuda/bin/compute-sanitizer
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
$CS --version | head -2
timeout 600 $CS --tool racecheck --print-level info python -X faulthandler tools/graph_san_min.py --only=c1 > $O/rcp_c1_graph.txt 2>&1; echo "rc c1 graph rc=$?"; tail -5 $O/rcp_c1_graph.txt
MAS_NO_GRAPH=1 timeout 600 $CS --tool racecheck python tools/graph_san_min.py --only=c1 > $O/rcp_c1_host.txt 2>&1; echo "rc c1 host rc=$?"; tail -2 $O/rcp_c1_host.txt
timeout 600 $CS --tool racecheck --racecheck-memcpy-async no python -X faulthandler tools/graph_san_min.py --only=c1 > $O/rcp_c1_graph_nomca.txt 2>&1; echo "rc c1 graph no-memcpy-async rc=$?"; tail -3 $O/rcp_c1_graph_nomca.txt
timeout 600 $CS --tool synccheck python -X faulthandler tools/graph_san_min.py --only=aniso > $O/rcp_sc_aniso_graph.txt 2>&1; echo "sc aniso graph rc=$?"; tail -4 $O/rcp_sc_aniso_graph.txt
