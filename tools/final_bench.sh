#!/bin/bash
# Round-end measurements on one B200: bench lines for every config + the C5 launch list.
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out
TAG=${1:-final}
timeout 900 python bench.py > gpurun_out/${TAG}_C5.log 2>&1
for c in C3 C4 C2 X1 X2; do
  timeout 600 python bench.py --config $c --no-cpu > gpurun_out/${TAG}_$c.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_ncu_launches_c5.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu \
  > gpurun_out/${TAG}_ncu_launches_c5.log 2>&1
timeout 600 python bench.py --config C3 --n-guides 10000 --no-cpu --no-e2e --steps 3 > gpurun_out/${TAG}_C3_10k.log 2>&1
timeout 600 python bench.py --config C3 --bulge 1,1 --no-cpu --no-e2e --steps 3 > gpurun_out/${TAG}_C3_bulge.log 2>&1
timeout 600 python bench.py --config C2 --bulge 2,2 --no-cpu --no-e2e --steps 5 > gpurun_out/${TAG}_C2_bulge.log 2>&1
