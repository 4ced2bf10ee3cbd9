# round 2, call 65: many-block geometry, survivors carried over 3 batches
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r65
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for i in 1 2; do
COF_LIB=$PWD/paper_conf_socc_jinv23_b200/libcofvK3.so timeout 300 python bench.py --config C5 $B > gpurun_out/r65/C5_K3_$i.jsonl 2> gpurun_out/r65/C5_K3_$i.err
timeout 300 python bench.py --config C5 $B > gpurun_out/r65/C5_K2_$i.jsonl 2> gpurun_out/r65/C5_K2_$i.err
done
