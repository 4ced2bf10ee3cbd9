# round 2, call 40 (and 45): checkpoint -- full GPU suite, full bench lines (all configs), C5 launch list,
# ncu --set full of the C5 single-pass kernel
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r40
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r40/smi.txt
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r40/gpu_tests.log 2>&1
timeout 900 python bench.py > gpurun_out/r40/C5.jsonl 2> gpurun_out/r40/C5.err
for c in C3 C4 C2 C1 X1 X2; do timeout 600 python bench.py --config $c --no-cpu --no-single-thread > gpurun_out/r40/$c.jsonl 2> gpurun_out/r40/$c.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r40/ref.jsonl 2> gpurun_out/r40/ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r40/ncu_launches_c5.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-fasta --no-single-thread \
  > gpurun_out/r40/ncu_launches_c5.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/r40/prof_C5 \
  python bench.py --config C5 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r40/prof_C5.log 2>&1
