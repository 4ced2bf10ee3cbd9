# round 2, call 69: many-block geometry variants on C5 (one group per step; 24 warps)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r69
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
L=$PWD/paper_conf_socc_jinv23_b200
for v in G1 W24; do COF_LIB=$L/libcofv$v.so timeout 300 python bench.py --config C5 $B > gpurun_out/r69/C5_$v.jsonl 2> gpurun_out/r69/C5_$v.err; done
timeout 300 python bench.py --config C5 $B > gpurun_out/r69/C5_base.jsonl 2> gpurun_out/r69/C5_base.err
