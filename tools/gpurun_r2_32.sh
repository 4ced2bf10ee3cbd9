# round 2, call 32: one-pass finder counting the next tile before the current look-back
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r32
timeout 300 python tools/stress_finder.py > gpurun_out/r32/stress.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C4 C3; do timeout 300 python bench.py --config $c $B > gpurun_out/r32/$c.jsonl 2> gpurun_out/r32/$c.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_finder_scan -s 2 -c 1 -o gpurun_out/r32/prof_find_C4 \
  python bench.py --config C4 --steps 2 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r32/prof_find_C4.log 2>&1
