python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider > gpurun_out/t13.log 2>&1; tail -1 gpurun_out/t13.log; grep FAILED gpurun_out/t13.log | head
python scripts/shard_quality.py > gpurun_out/r2_shard_quality.txt 2>&1; cat gpurun_out/r2_shard_quality.txt | cut -c1-600
