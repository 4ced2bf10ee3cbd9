# round 2, call 63 (final: many-block geometry with 4-batch queues): checkpoint -- full GPU suite, full bench lines (all configs), C5 launch list,
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r63
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r63/smi.txt
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r63/gpu_tests.log 2>&1
timeout 900 python bench.py > gpurun_out/r63/C5.jsonl 2> gpurun_out/r63/C5.err
for c in C3 C4 C2 C1 X1 X2; do timeout 600 python bench.py --config $c --no-cpu --no-single-thread > gpurun_out/r63/$c.jsonl 2> gpurun_out/r63/$c.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r63/ref.jsonl 2> gpurun_out/r63/ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r63/ncu_launches_c5.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-fasta --no-single-thread \
  > gpurun_out/r63/ncu_launches_c5.log 2>&1
