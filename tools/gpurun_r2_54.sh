# round 2, call 54: ncu --set full of the final single pass on C4 (four words per lane) and C3
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r54
for c in C4 C3; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/r54/prof_$c \
  python bench.py --config $c --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r54/prof_$c.log 2>&1
done
