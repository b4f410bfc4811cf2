# A/B probe of V_MIDDLE segred on the n*m = 2^26 sweep (middle vs top/flat around the crossovers)
mkdir -p gpurun_out
timeout 300 python tools/version_probe.py 0 1 2 3 4 5 6 7 8 12 13 14 15 16 17 18 19 20 21 22 --ops segred --versions top,middle,flat > gpurun_out/ab_mid.json 2>&1; cat gpurun_out/ab_mid.json
