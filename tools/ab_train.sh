# segred MIDDLE vs FLAT around n = 8 at the tuner's training sizes (2^25, 2^27) and the test size
for L in 25 26 27; do timeout 200 python tools/version_probe.py 2 3 4 5 --ops segred --versions middle,flat --log2n $L; done
