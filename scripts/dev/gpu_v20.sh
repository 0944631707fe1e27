# the driver's multi-rank launch form at N=1 (torchrun, NCCL process group), both arms
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_v20.log 2>&1; echo build rc=$?
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 1 --steps 5 --warmup 3 > gpurun_out/bench_tr1.json 2> gpurun_out/bench_tr1.err; echo "torchrun ours rc=$?"; cut -c1-250 gpurun_out/bench_tr1.json
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29512 bench.py --impl reference --gpus 1 --steps 2 --warmup 1 > gpurun_out/bench_tr1_ref.json 2> gpurun_out/bench_tr1_ref.err; echo "torchrun ref rc=$?"; cut -c1-250 gpurun_out/bench_tr1_ref.json
