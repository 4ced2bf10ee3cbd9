# round 2, call 60: L > 32 PAM path only in the generic kernels (C4 regression check)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r60
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -x -q > gpurun_out/r60/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 X2 C3 C5; do timeout 300 python bench.py --config $c $B > gpurun_out/r60/$c.jsonl 2> gpurun_out/r60/$c.err; done
