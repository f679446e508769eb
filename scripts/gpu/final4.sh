TAG=r2s2c bash scripts/gpu/campaign_b.sh
( time python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/r2s2c_gputests.log 2>&1 ) 2> gpurun_out/r2s2c_gputests.time
tail -3 gpurun_out/r2s2c_gputests.log; cat gpurun_out/r2s2c_gputests.time
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
