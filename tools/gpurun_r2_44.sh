# round 2, call 44: two plane words per lane for dense PAMs (C3, C2 via COF_SPARSE=1; C5 via variant)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r44
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C3 C2; do
  timeout 300 python bench.py --config $c $B > gpurun_out/r44/$c.jsonl 2> gpurun_out/r44/$c.err
  COF_SPARSE=1 timeout 300 python bench.py --config $c $B > gpurun_out/r44/${c}_w2.jsonl 2> gpurun_out/r44/${c}_w2.err
done
timeout 300 python bench.py --config C5 $B > gpurun_out/r44/C5.jsonl 2> gpurun_out/r44/C5.err
COF_LIB=$PWD/paper_conf_socc_jinv23_b200/libcofM2.so timeout 300 python bench.py --config C5 $B > gpurun_out/r44/C5_w2.jsonl 2> gpurun_out/r44/C5_w2.err
