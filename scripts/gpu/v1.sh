set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
( time python -m pytest tests -q -m gpu -p no:cacheprovider --durations=25 > gpurun_out/v1_gputests.log 2>&1 ) 2> gpurun_out/v1_gputests.time
tail -3 gpurun_out/v1_gputests.log
python bench.py > gpurun_out/v1_bench.json 2> gpurun_out/v1_bench.err
tail -c 3000 gpurun_out/v1_bench.json
