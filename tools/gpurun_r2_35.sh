# round 2, call 35: survivors carried over up to K batches (few-block plans), + C4/C3 profiles
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r35
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
L=paper_conf_socc_jinv23_b200
for c in C3 C4; do timeout 300 python bench.py --config $c $B > gpurun_out/r35/base_$c.jsonl 2> gpurun_out/r35/base_$c.err; done
for v in K2 K3; do for c in C3 C4; do
  COF_LIB=$L/libcofvar$v.so timeout 300 python bench.py --config $c $B > gpurun_out/r35/${v}_$c.jsonl 2> gpurun_out/r35/${v}_$c.err; done; done
for c in C4 C3; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/r35/prof_$c \
  python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r35/prof_$c.log 2>&1
done
