# round 2, call 30: one-pass finder with 65536-start tiles and a 256-tile look-back window
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r30
timeout 300 python tools/stress_finder.py > gpurun_out/r30/stress.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 C3; do timeout 300 python bench.py --config $c $B > gpurun_out/r30/$c.jsonl 2> gpurun_out/r30/$c.err; done
for c in C4; do COF_PATH=twocall timeout 600 python bench.py --config $c $B > gpurun_out/r30/${c}_twocall.jsonl 2> gpurun_out/r30/${c}_twocall.err; done
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r30/tests.log 2>&1
