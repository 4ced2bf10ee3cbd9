# round 2, call 43: 4 plane words per lane for sparse PAMs (variant library)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r43
L=$PWD/paper_conf_socc_jinv23_b200/libcofW4.so
COF_LIB=$L COF_SPARSE=1 timeout 900 python -m pytest tests/test_gpu_single.py -x -q > gpurun_out/r43/tests_w4.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
COF_LIB=$L timeout 300 python bench.py --config C4 $B > gpurun_out/r43/C4_W4.jsonl 2> gpurun_out/r43/C4_W4.err
timeout 300 python bench.py --config C4 $B > gpurun_out/r43/C4.jsonl 2> gpurun_out/r43/C4.err
