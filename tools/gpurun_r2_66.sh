# round 2, call 66: final -- many-block survivors over 3 batches; tests, C5 default bench line
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r66
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r66/gpu_tests.log 2>&1
timeout 900 python bench.py > gpurun_out/r66/C5.jsonl 2> gpurun_out/r66/C5.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r66/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r66/smoke.log
