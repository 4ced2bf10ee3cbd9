# round 2, call 13: full GPU suite on the single-pass default + C4 profile + full C5 bench line
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r2_t13_all.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof13_C4 python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > /dev/null 2>&1
timeout 900 python bench.py --config C5 > gpurun_out/r2_b13_C5_full.jsonl 2> gpurun_out/r2_b13_C5_full.err
timeout 900 python bench.py --config C3 --no-cpu --no-single-thread > gpurun_out/r2_b13_C3_full.jsonl 2> gpurun_out/r2_b13_C3_full.err
