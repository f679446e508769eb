TAG=${TAG:-r2s2b}
for c in web_40m_2200m sbm_1m_20m rmat_4m_70m road_50m_110m kmer_171m_360m; do
  python bench.py --config $c > gpurun_out/${TAG}_bench_$c.json 2> gpurun_out/${TAG}_bench_$c.err
  tail -c 300 gpurun_out/${TAG}_bench_$c.err
done
