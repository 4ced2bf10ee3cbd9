# round 2, call 56: N=2 bench (two ranks sharing one GPU over gloo) at full size, C5 and C3
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/r56
df -h /dev/shm > gpurun_out/r56/shm.txt
for c in C5 C3; do
COF_DIST_BACKEND=gloo timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29561 bench.py --gpus 2 --config $c --steps 3 --warmup 3 > gpurun_out/r56/${c}_n2.jsonl 2> gpurun_out/r56/${c}_n2.err
done
