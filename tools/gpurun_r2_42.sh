# round 2, call 42: words-per-lane generalisation; sparse PAMs (Cas12a) take 2 plane words per lane
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r42
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -x -q > gpurun_out/r42/tests.log 2>&1
COF_SPARSE=1 timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -x -q > gpurun_out/r42/tests_sparse.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
L=paper_conf_socc_jinv23_b200
for c in C4 C3 C5 C2; do timeout 300 python bench.py --config $c $B > gpurun_out/r42/$c.jsonl 2> gpurun_out/r42/$c.err; done
COF_SPARSE=0 timeout 300 python bench.py --config C4 $B > gpurun_out/r42/C4_nosparse.jsonl 2> gpurun_out/r42/C4_nosparse.err
COF_LIB=$L/libcof_W4.so timeout 300 python bench.py --config C4 $B > gpurun_out/r42/C4_W4.jsonl 2> gpurun_out/r42/C4_W4.err
