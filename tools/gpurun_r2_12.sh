# round 2, call 12: two kernel geometries in one library (few: 20 warps x 2 sites, many: 28 x 1),
# one-survivor-per-entry verification rounds with re-append, sleeping tile wait
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_resident.py -x -q 2>&1 | tail -3 > gpurun_out/r2_t12_single.log
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C5 C3 C4 C2 C1; do timeout 600 python bench.py --config $c $B > gpurun_out/r2_b12_${c}.jsonl 2> gpurun_out/r2_b12_${c}.err; done
COF_PATH=fused timeout 600 python bench.py --config C3 $B > gpurun_out/r2_b12_fused_C3.jsonl 2> gpurun_out/r2_b12_fused_C3.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof12_C5 python bench.py --config C5 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof12_C3 python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
