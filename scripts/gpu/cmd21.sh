python -m pytest tests/test_gpu_parity.py -q -p no:cacheprovider -x > gpurun_out/t18.log 2>&1; tail -3 gpurun_out/t18.log
python scripts/exp_device_loop.py 2>&1 | tail -8
