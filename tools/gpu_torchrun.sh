cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --steps 20 --warmup 3 --no-cpu --e2e-steps 5 > gpurun_out/torchrun1.json 2> gpurun_out/torchrun1.err; echo "exit $?" >> gpurun_out/torchrun1.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 bench.py --gpus 2 --steps 20 --warmup 3 --no-e2e --payload-mib 16 > gpurun_out/torchrun2.json 2> gpurun_out/torchrun2.err; echo "exit $?" >> gpurun_out/torchrun2.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/ref.json 2> gpurun_out/ref.err; echo "exit $?" >> gpurun_out/ref.err
