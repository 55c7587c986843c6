for a in "140 23 1" "67 9 2" "200 5 2" "130 7 3"; do python tools/cg_dump.py $a 2>/dev/null | tail -1; done > gpurun_out/dump9.log
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/check3_tests.log 2>&1; tail -n 2 gpurun_out/check3_tests.log
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29535 bench.py --impl reference --gpus 2 --steps 3 --warmup 3 2>/dev/null | tail -1 > gpurun_out/mr_ref2.log
