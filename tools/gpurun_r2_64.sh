# round 2, call 64: checks build on the final many-block geometry (C5 full size, single-pass tests)
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r64
CL=$PWD/paper_conf_socc_jinv23_b200/libcofchecks.so
COF_LIB=$CL timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -q > gpurun_out/r64/checks_tests.log 2>&1
COF_LIB=$CL timeout 600 python bench.py --config C5 --steps 2 --warmup 3 --no-cpu --no-single-thread --no-fasta > gpurun_out/r64/checks_C5.jsonl 2> gpurun_out/r64/checks_C5.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r64/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r64/smoke.log
