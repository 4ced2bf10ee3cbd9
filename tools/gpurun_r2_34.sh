# round 2, call 34: GPU tests and full-size configs against the COF_CHECKS build (device-side
# invariant traps; compute-sanitizer is closed on this pool), then the product build's tests
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r34
CL=$PWD/paper_conf_socc_jinv23_b200/libcofchecks.so
COF_LIB=$CL timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r34/checks_tests.log 2>&1
COF_LIB=$CL timeout 600 python tools/sanitize_cases.py > gpurun_out/r34/checks_cases.log 2>&1; echo "rc=$?" >> gpurun_out/r34/checks_cases.log
for c in C5 C3 C4 C2 C1; do COF_LIB=$CL timeout 600 python bench.py --config $c --steps 2 --warmup 3 --no-cpu --no-single-thread --no-fasta > gpurun_out/r34/checks_$c.jsonl 2> gpurun_out/r34/checks_$c.err; done
