# round 2, call 39: search_host finishes every completed chunk at once (D2H not delayed)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r39
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi.py -x -q > gpurun_out/r39/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta"
for c in C3 C5 C4; do timeout 600 python bench.py --config $c $B > gpurun_out/r39/$c.jsonl 2> gpurun_out/r39/$c.err; done
for c in C3 C5; do COF_REC_BUFS=2 COF_PLANE_BUFS=2 timeout 600 python bench.py --config $c $B > gpurun_out/r39/${c}_2buf.jsonl 2> gpurun_out/r39/${c}_2buf.err; done
