# round 2, call 37: branch-free verification rounds (fail masks stored), search_host without a
# per-chunk host sync (counts read one chunk late, restart on overflow), split fill measured again
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r37
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r37/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta"
for c in C3 C5 C4; do timeout 600 python bench.py --config $c $B > gpurun_out/r37/$c.jsonl 2> gpurun_out/r37/$c.err; done
for c in C3 C5; do COF_SPLIT_FILL=1 COF_TRACE=1 timeout 600 python bench.py --config $c $B > gpurun_out/r37/${c}_split.jsonl 2> gpurun_out/r37/${c}_split.err; done
