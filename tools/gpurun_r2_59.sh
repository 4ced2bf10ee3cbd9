# round 2, call 59: single pass for L > 32 when the compared span fits one word (X2-like shapes)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r59
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r59/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta"
for c in X2 C5 C3 C4; do timeout 300 python bench.py --config $c $B > gpurun_out/r59/$c.jsonl 2> gpurun_out/r59/$c.err; done
