( time python -m pytest tests -q -m gpu -p no:cacheprovider > gpurun_out/r2s2e_gputests.log 2>&1 ) 2> gpurun_out/r2s2e_gputests.time
tail -2 gpurun_out/r2s2e_gputests.log; tail -3 gpurun_out/r2s2e_gputests.time
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
python bench.py > gpurun_out/r2s2e_bench_web_40m_2200m.json 2> gpurun_out/r2s2e_bench.err
tail -c 700 gpurun_out/r2s2e_bench_web_40m_2200m.json
