timeout 300 python tools/timeline.py 8192 1024 dev 20
timeout 300 python tools/timeline.py 8192 512 dev 20
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --virtual-slots 1 --steps 2 --warmup 3 --no-cpu > gpurun_out/mp_bench.json 2> gpurun_out/mp_bench.err; echo "torchrun rc=$?"; tail -c 600 gpurun_out/mp_bench.json
