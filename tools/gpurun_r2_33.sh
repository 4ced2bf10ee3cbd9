# round 2, call 33: one-pass finder tile size sweep (words per thread 8 / 4 / 2)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r33
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
L=paper_conf_socc_jinv23_b200
for v in S4 S2; do for c in C4 C3; do
  COF_LIB=$L/libcof_$v.so timeout 300 python bench.py --config $c $B > gpurun_out/r33/${v}_$c.jsonl 2> gpurun_out/r33/${v}_$c.err; done; done
