# round 2, call 27: geometry sweep of the single pass (variant libraries via COF_LIB)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r27
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
L=paper_conf_socc_jinv23_b200
for c in C3 C4 C5; do timeout 600 python bench.py --config $c $B > gpurun_out/r27/base_$c.jsonl 2> gpurun_out/r27/base_$c.err; done
for v in F1 F2 F3; do for c in C3 C4; do
  COF_LIB=$L/libcof_$v.so timeout 600 python bench.py --config $c $B > gpurun_out/r27/${v}_$c.jsonl 2> gpurun_out/r27/${v}_$c.err; done; done
for v in M1 M2 M3; do
  COF_LIB=$L/libcof_$v.so timeout 600 python bench.py --config C5 $B > gpurun_out/r27/${v}_C5.jsonl 2> gpurun_out/r27/${v}_C5.err; done
