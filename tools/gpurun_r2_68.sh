# round 2, call 68: ncu --set full of the final single pass on C5 (many-block geometry, 4-batch queues)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r68
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/r68/prof_C5 \
  python bench.py --config C5 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r68/prof_C5.log 2>&1
