#!/bin/bash
# ncu captures of the C3 hot kernels (run on the GPU box; reports stay in /tmp, text
# summaries go to gpurun_out/).  Usage: bash tools/prof_c3.sh [CONFIG] [TAG]
export PATH=/usr/local/cuda/bin:$PATH
CFG=${1:-C3}; TAG=${2:-c3}
P=/tmp/prof; mkdir -p $P gpurun_out
B="python bench.py --config $CFG --steps 1 --warmup 1 --no-e2e --no-cpu"
NCU="ncu --set full --clock-control none --import-source on -f"
timeout 400 $NCU -k regex:cof_comparer -c 1 -o $P/${TAG}_cmp $B > gpurun_out/ncu_${TAG}_cmp.log 2>&1
timeout 400 $NCU -k regex:cof_finder -c 1 -o $P/${TAG}_find $B > gpurun_out/ncu_${TAG}_find.log 2>&1
COF_FUSED=1 timeout 400 $NCU -k regex:cof_comparer_fused -c 1 -o $P/${TAG}f_cmp $B > gpurun_out/ncu_${TAG}f_cmp.log 2>&1
for r in $P/*.ncu-rep; do
  b=$(basename $r .ncu-rep)
  python tools/ncu_hot.py $r 40 > gpurun_out/$b.hot.txt 2>&1
  ncu -i $r --page details > gpurun_out/$b.details.txt 2>&1
done
