# round 2, call 49: ncu --set full of the search kernel (cof_find_pam item lists) on C4 and C3
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r49
for c in C4 C3; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_finder_kernel -s 1 -c 1 -o gpurun_out/r49/prof_find_$c \
  python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r49/prof_find_$c.log 2>&1
done
