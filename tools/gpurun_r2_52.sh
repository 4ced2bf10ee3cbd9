# round 2, call 52: finder pass 2 bit index with one FLO; 4 plane words per lane for sparse PAMs
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r52
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "pam or capacity or random_small or configs" > gpurun_out/r52/tests.log 2>&1
COF_LIB=$PWD/paper_conf_socc_jinv23_b200/libcofW4.so COF_SPARSE=1 timeout 900 python -m pytest tests/test_gpu_single.py -x -q > gpurun_out/r52/tests_w4.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 C3; do timeout 300 python bench.py --config $c $B > gpurun_out/r52/$c.jsonl 2> gpurun_out/r52/$c.err; done
for i in 1 2; do COF_LIB=$PWD/paper_conf_socc_jinv23_b200/libcofW4.so timeout 300 python bench.py --config C4 $B > gpurun_out/r52/C4_W4_$i.jsonl 2> gpurun_out/r52/C4_W4_$i.err; timeout 300 python bench.py --config C4 $B > gpurun_out/r52/C4_W2_$i.jsonl 2> gpurun_out/r52/C4_W2_$i.err; done
