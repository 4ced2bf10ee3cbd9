# round 2, call 67: few-block configs on the many-block geometry (COF_FEW_MAXB=0)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r67
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C3 C4 C2; do
COF_LIB=$PWD/paper_conf_socc_jinv23_b200/libcofvM.so timeout 300 python bench.py --config $c $B > gpurun_out/r67/${c}_many.jsonl 2> gpurun_out/r67/${c}_many.err
timeout 300 python bench.py --config $c $B > gpurun_out/r67/${c}.jsonl 2> gpurun_out/r67/${c}.err
done
