set -x
timeout 1200 ncu --set full --import-source on --clock-control none --kernel-name-base mangled -k regex:k_warpILb0ELb1ELi512 -c 2 -f -o gpurun_out/r2s2_kwarp_full python scripts/profile_run.py --runs 1 > gpurun_out/r2s2_kwarp_full.log 2>&1
ls -la gpurun_out/
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 1 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 1 --distributed --steps 5 --warmup 3 > gpurun_out/r2s2_dist1.json 2> gpurun_out/r2s2_dist1.err
tail -c 1500 gpurun_out/r2s2_dist1.json
SHARDS=1,2,4,8 timeout 1200 python scripts/shard_quality.py > gpurun_out/r2s2_shard_quality.txt 2>&1
cut -c1-300 gpurun_out/r2s2_shard_quality.txt
