mkdir -p gpurun_out
for c in road rmat er; do timeout 600 python tools/sweep.py --config $c --sources 6 --profile --sets '[{}]' > gpurun_out/sw5_$c.log 2>&1; done
for c in road rmat er; do timeout 300 python tools/trace.py --config $c --rows 40 > gpurun_out/trace5_$c.log 2>&1; done
timeout 900 python -m pytest tests -m gpu -x -q -k "perturbation or trace or controller" > gpurun_out/pytest5.log 2>&1; echo pytest=$? >> gpurun_out/pytest5.log
