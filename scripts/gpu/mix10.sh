for v in cur v84 cur v84; do NULPA_LIB=libs_ab/libnulpa_$v.so CONFIG=kmer_171m_360m PSETS="kmer_$v:" bash scripts/gpu/ab_params.sh; done
