mkdir -p gpurun_out
for lib in libsplit_ga.so libsplit_ga_b2.so; do
  echo "== $lib"
  export SPLIT_LIB=paper_conf_icpp_luoyww0023_b200/lib/$lib
  python tools/ga_c2_probe.py 2>&1 | tail -1
  python tools/ga_big_probe.py 2>&1 | tail -4
done
SPLIT_LIB=paper_conf_icpp_luoyww0023_b200/lib/libsplit_ga_b2.so timeout 900 python -m pytest tests/test_gpu_ga.py -q -x -p no:cacheprovider -k "c2_full_size_first or large_population or hbm_regime or eight_large or local_islands or c1_trajectory" 2>&1 | tail -2
