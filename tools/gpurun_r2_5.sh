# round 2, call 5: single pass v4 (hand-reduced filter circuits, two-step survivor verification,
# count-bounded append loop) + the masks path for comparison
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests/test_gpu_single.py -x -q 2>&1 | tail -5 > gpurun_out/r2_t5_single.log
for c in C5 C3 C4 C2; do timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e > gpurun_out/r2_b5_$c.jsonl 2> gpurun_out/r2_b5_$c.err; done
for c in C5 C3 C4; do COF_PATH=fused timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e > gpurun_out/r2_b5f_$c.jsonl 2> gpurun_out/r2_b5f_$c.err; done
COF_PATH=twocall timeout 600 python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e > gpurun_out/r2_b5t_C4.jsonl 2> gpurun_out/r2_b5t_C4.err
for c in C3 C5; do timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/prof5_single_$c python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/prof5_single_$c.log 2>&1; done
