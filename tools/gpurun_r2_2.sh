# round 2, call 2: single-pass kernel parity + first bench lines
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -30 > gpurun_out/r2_t2_single.log
timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "full_size or configs_scaled or uniform or worked or c1_full" 2>&1 | tail -30 > gpurun_out/r2_t2_parity.log
for c in C5 C3 C4 C2; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta > gpurun_out/r2_b2_$c.jsonl 2> gpurun_out/r2_b2_$c.err; done
tail -3 gpurun_out/r2_t2_single.log gpurun_out/r2_t2_parity.log
