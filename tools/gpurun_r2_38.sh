# round 2, call 38: search_host with 3 plane sets, 3 record buffers (counts read two chunks
# late), split fill by default
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r38
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multi.py tests/test_cli.py -x -q > gpurun_out/r38/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta"
for c in C3 C5 C4; do COF_TRACE=1 timeout 600 python bench.py --config $c $B > gpurun_out/r38/$c.jsonl 2> gpurun_out/r38/$c.err; done
for c in C3 C5; do COF_SPLIT_FILL=0 timeout 600 python bench.py --config $c $B > gpurun_out/r38/${c}_nosplit.jsonl 2> gpurun_out/r38/${c}_nosplit.err; done
