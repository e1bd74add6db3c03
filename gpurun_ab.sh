set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -5
for lib in paper_conf_ppopp_wangfl21_b200/libsssp.so ab/libsssp_noca.so; do
  echo "== $lib"
  for c in road rmat er; do
    SSSP_LIB=$lib timeout 300 python tools/sweep.py --config $c --sources 3 --sets '[{}]' --deltas "$( [ $c = road ] && echo 12 || ([ $c = rmat ] && echo 3 || echo 15))"
  done
done
