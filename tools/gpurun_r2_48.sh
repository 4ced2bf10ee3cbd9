# round 2, call 48: CUDA-graph replay of launch-bound bench steps (C1, C2, X1, X2)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r48
timeout 900 python -m pytest tests/test_gpu_bench.py -x -q > gpurun_out/r48/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C2 C1 X1 X2 C4; do timeout 300 python bench.py --config $c $B > gpurun_out/r48/$c.jsonl 2> gpurun_out/r48/$c.err; done
COF_GRAPH=0 timeout 300 python bench.py --config C2 $B > gpurun_out/r48/C2_eager.jsonl 2> gpurun_out/r48/C2_eager.err
