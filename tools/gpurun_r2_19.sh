# round 2, call 19: merged-strand append only for sparse PAMs
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_resident.py -x -q 2>&1 | tail -2 > gpurun_out/r2_t19_single.log
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C3 C4 C2 C5 C1; do timeout 600 python bench.py --config $c $B > gpurun_out/r2_b19_${c}.jsonl 2> gpurun_out/r2_b19_${c}.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof19_C4 python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof19_C3 python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
