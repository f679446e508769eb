( time python -m pytest tests -q -m gpu -p no:cacheprovider --durations=15 > gpurun_out/r2s2_gputests.log 2>&1 ) 2> gpurun_out/r2s2_gputests.time
tail -22 gpurun_out/r2s2_gputests.log; cat gpurun_out/r2s2_gputests.time
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
