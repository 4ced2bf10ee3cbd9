# round 2, call 26: filter tables without N entries (N read as A), no valid-mask for uniform
# thresholds, two groups per filter step for many-block plans (immediate table offsets)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r26
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -x -q > gpurun_out/r26/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C5 C3 C4 C2; do timeout 600 python bench.py --config $c $B > gpurun_out/r26/$c.jsonl 2> gpurun_out/r26/$c.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/r26/prof_C5 \
  python bench.py --config C5 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r26/prof_C5.log 2>&1
