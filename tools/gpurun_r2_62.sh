# round 2, call 62: many-block geometry with a 2-stage ring and 4-batch queues (survivors
# carried over 1 or 2 batches)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r62
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
L=$PWD/paper_conf_socc_jinv23_b200
COF_LIB=$L/libcofvA.so COF_SINGLE=1 timeout 600 python -m pytest tests/test_gpu_single.py -x -q > gpurun_out/r62/tests_A.log 2>&1
for v in A B; do COF_LIB=$L/libcofv$v.so timeout 300 python bench.py --config C5 $B > gpurun_out/r62/C5_$v.jsonl 2> gpurun_out/r62/C5_$v.err; done
timeout 300 python bench.py --config C5 $B > gpurun_out/r62/C5_base.jsonl 2> gpurun_out/r62/C5_base.err
