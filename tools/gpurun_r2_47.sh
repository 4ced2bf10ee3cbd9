# round 2, call 47: final code -- smoke(), GPU suite against the COF_CHECKS build (also with the
# sparse geometry forced), checks build on the full-size configs
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r47
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r47/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r47/smoke.log
CL=$PWD/paper_conf_socc_jinv23_b200/libcofchecks.so
COF_LIB=$CL timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r47/checks_tests.log 2>&1
COF_LIB=$CL COF_SPARSE=1 timeout 900 python -m pytest tests/test_gpu_single.py tests/test_gpu_parity.py -q > gpurun_out/r47/checks_tests_sparse.log 2>&1
COF_LIB=$CL timeout 600 python tools/sanitize_cases.py > gpurun_out/r47/checks_cases.log 2>&1; echo "rc=$?" >> gpurun_out/r47/checks_cases.log
for c in C5 C3 C4; do COF_LIB=$CL timeout 600 python bench.py --config $c --steps 2 --warmup 3 --no-cpu --no-single-thread --no-fasta > gpurun_out/r47/checks_$c.jsonl 2> gpurun_out/r47/checks_$c.err; done
