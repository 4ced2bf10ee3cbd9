# round 2, call 51: PAM letter count as a template parameter of the single pass (2 / 4 letters)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r51
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -x -q > gpurun_out/r51/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 C3 C5 C2; do timeout 300 python bench.py --config $c $B > gpurun_out/r51/$c.jsonl 2> gpurun_out/r51/$c.err; done
