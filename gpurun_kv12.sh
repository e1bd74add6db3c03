timeout 500 python tools/sweep.py --config road --sources 6 --profile --sets '[{"delta_init": 4096}, {"delta_init": 4096, "delta_mode": 1}]' 2>&1 | grep kernel_ms
