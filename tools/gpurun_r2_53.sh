# round 2, call 53 (final): checkpoint -- full GPU suite, full bench lines (all configs), C5 launch list,
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r53
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/r53/smi.txt
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r53/gpu_tests.log 2>&1
timeout 900 python bench.py > gpurun_out/r53/C5.jsonl 2> gpurun_out/r53/C5.err
for c in C3 C4 C2 C1 X1 X2; do timeout 600 python bench.py --config $c --no-cpu --no-single-thread > gpurun_out/r53/$c.jsonl 2> gpurun_out/r53/$c.err; done
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/r53/ref.jsonl 2> gpurun_out/r53/ref.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/r53/ncu_launches_c5.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu --no-fasta --no-single-thread \
  > gpurun_out/r53/ncu_launches_c5.log 2>&1
CL=$PWD/paper_conf_socc_jinv23_b200/libcofchecks.so
COF_LIB=$CL COF_SPARSE=1 timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -q > gpurun_out/r53/checks_tests_sparse.log 2>&1
COF_LIB=$CL timeout 600 python bench.py --config C4 --steps 2 --warmup 3 --no-cpu --no-single-thread --no-fasta > gpurun_out/r53/checks_C4.jsonl 2> gpurun_out/r53/checks_C4.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r53/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r53/smoke.log
