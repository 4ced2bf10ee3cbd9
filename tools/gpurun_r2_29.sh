# round 2, call 29: one-pass finder, next ticket drawn after the current tile's count
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r29
timeout 300 python -m pytest tests/test_gpu_multi.py -k busy_stream -x -q > gpurun_out/r29/busy.log 2>&1
timeout 300 python -m pytest tests/test_gpu_parity.py -k "pam or capacity" -x -q > gpurun_out/r29/pam.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 C3; do timeout 300 python bench.py --config $c $B > gpurun_out/r29/$c.jsonl 2> gpurun_out/r29/$c.err; done
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r29/tests.log 2>&1
