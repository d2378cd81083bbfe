#!/bin/bash
# where k_aniso's DRAM reads come from: L2 read sectors (all sources / from
# L1TEX = plain loads), their misses, DRAM bytes; PCGA and APPLY launches
cd "$(dirname "$0")/.."
O=gpurun_out; TAG=${TAG:-r3b}
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1 || exit 1
M=dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_op_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_op_read_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_read_lookup_miss.sum,lts__t_sectors_op_write.sum,gpu__time_duration.sum
for skip in 0 1 2 3; do
  MAS_NO_GRAPH=1 /usr/local/cuda/bin/ncu --metrics $M --clock-control none -k regex:k_aniso --launch-skip $skip --launch-count 1 --csv \
    python tools/prof_driver.py --config C2a > $O/${TAG}_traffic_$skip.csv 2>/dev/null
  echo "== launch $skip"; grep -E "k_aniso" $O/${TAG}_traffic_$skip.csv | awk -F'","' '{print $5" | "$(NF-2)" "$(NF-1)" "$NF}' | head -12
done
