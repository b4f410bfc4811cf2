# A/B of experiment builds of the flat engine (run under gpurun):
#   LIBS="libifl.so libifl_x.so" SHAPES="1 64 ..." TESTLIB=libifl_x.so bash tools/ab_scan.sh
L=$PWD/paper_conf_ppopp_henriksenteo19_b200
for lib in ${TESTLIBS:-libifl.so}; do
  IFL_LIB_PATH=$L/$lib timeout 300 python -m pytest tests -m gpu -q -x -k "scan or seeded" 2>&1 | tail -1
done
for lib in ${LIBS:-libifl.so}; do
  IFL_LIB_PATH=$L/$lib timeout 120 python tools/flat_probe.py ${SHAPES:-1 64 1024 8192 65536 262144}
done
