# Experiment variant of flat.cu only: bash tools/vbuild.sh TAG "-DX=1 -DY=2"
IFL_BUILD_TAG=$1 IFL_BUILD_EXTRA="$2" IFL_BUILD_ONLY="${3:-flat.cu}" python -m paper_conf_ppopp_henriksenteo19_b200.build | tail -1
