#!/bin/bash
# narrowing the synccheck / racecheck failures of round-2 graph_sanitize.sh
cd "$(dirname "$0")/.."
out=gpurun_out; mkdir -p $out
CS=/usr/local/cuda/bin/compute-sanitizer
python -c "import __graft_entry__ as g; g.build()" || exit 1
nvcc -gencode arch=compute_100a,code=sm_100a -o tools/graph_cond_check tools/graph_cond_check.cu
run() { # name, env, tool, args
  local name=$1 envs=$2 tool=$3; shift 3
  env $envs timeout 600 $CS --tool $tool --print-limit 20 "$@" > $out/san2_$name.txt 2>&1
  echo "$name rc=$?: $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|Program hit|Error:' $out/san2_$name.txt | head -2 | tr '\n' ' ')"
}
run rc_repro "" racecheck tools/graph_cond_check
run sc_repro "" synccheck tools/graph_cond_check
run rc_c1_graph "" racecheck python tools/graph_san_min.py --only=c1
run rc_c1_nograph "MAS_NO_GRAPH=1" racecheck python tools/graph_san_min.py --only=c1
run rc_all_nograph "MAS_NO_GRAPH=1" racecheck python tools/graph_san_min.py
run sc_aniso_graph "" synccheck python tools/graph_san_min.py --only=aniso
run sc_aniso_nograph "MAS_NO_GRAPH=1" synccheck python tools/graph_san_min.py --only=aniso
run sc_p2p_graph "" synccheck python tools/graph_san_min.py --only=p2p
run mc_aniso_nograph "MAS_NO_GRAPH=1" memcheck python tools/graph_san_min.py --only=aniso,p2p
