set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
df -h /dev/shm | tail -1
python -m pytest tests -m gpu -x -q -k "multi or bench or grid_exchange" 2>&1 | tail -30 > gpurun_out/r2_t1_multi.log
python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/r2_t1_all.log
python bench.py --config C5 --steps 10 --warmup 3 > gpurun_out/r2_b1_c5.jsonl 2> gpurun_out/r2_b1_c5.err
python bench.py --config C3 --steps 10 --warmup 3 --no-cpu --no-single-thread > gpurun_out/r2_b1_c3.jsonl 2> gpurun_out/r2_b1_c3.err
python bench.py --config C4 --steps 10 --warmup 3 --no-cpu --no-single-thread > gpurun_out/r2_b1_c4.jsonl 2> gpurun_out/r2_b1_c4.err
tail -3 gpurun_out/r2_t1_multi.log gpurun_out/r2_t1_all.log
