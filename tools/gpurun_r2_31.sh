# round 2, call 31: ncu of the one-pass finder (C4)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r31
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_finder_scan -s 2 -c 1 -o gpurun_out/r31/prof_find_C4 \
  python bench.py --config C4 --steps 2 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r31/prof_find_C4.log 2>&1
