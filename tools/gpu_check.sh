set -x
nvidia-smi -L
timeout 900 python -m pytest tests/test_ipc_group.py -x -q 2>&1 | tail -15
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 5 --warmup 3 --transport p2p --config cfg3a_schnakenberg_2m 2>&1 | tail -3
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 1 --steps 5 --warmup 3 --transport nccl --config cfg3a_schnakenberg_2m 2>&1 | tail -3
