# round 2, call 8: single pass v7 (one flush site, drain pass) + 20-warp variant (COF_LIB)
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -3 > gpurun_out/r2_t8_single.log
for c in C5 C3 C4; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e > gpurun_out/r2_b8_$c.jsonl 2> gpurun_out/r2_b8_$c.err; done
for c in C5 C3 C4; do COF_LIB=$PWD/variants/libcof_sw20.so timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e > gpurun_out/r2_b8w_$c.jsonl 2> gpurun_out/r2_b8w_$c.err; done
COF_LIB=$PWD/variants/libcof_sw20.so timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -3 > gpurun_out/r2_t8w_single.log
for c in C3 C5; do timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof8_single_$c python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/prof8_single_$c.log 2>&1; done
