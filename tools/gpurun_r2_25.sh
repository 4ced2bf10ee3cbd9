# round 2, call 25: single pass with direct per-lane queue appends (no owner list), 4-batch queue
# for few-block plans, survivor append predicate instead of per-block masking
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r25
timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -x -q > gpurun_out/r25/tests.log 2>&1
B="--steps 10 --warmup 3 --no-cpu --no-single-thread --no-fasta --no-e2e"
for c in C3 C4 C5 C2; do timeout 600 python bench.py --config $c $B > gpurun_out/r25/$c.jsonl 2> gpurun_out/r25/$c.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cof_single -s 1 -c 1 -o gpurun_out/r25/prof_C3 \
  python bench.py --config C3 --steps 1 --warmup 3 --no-e2e --no-cpu --no-fasta --no-single-thread > gpurun_out/r25/prof_C3.log 2>&1
