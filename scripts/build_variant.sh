#!/bin/bash
# usage: scripts/build_variant.sh NAME "-DFLAG=V ..."  -> variants/libopp_NAME.so (measurement A/B builds)
mkdir -p variants
OPP_NVCC_EXTRA="$2" OPP_LIB_OUT=$PWD/variants/libopp_$1.so python -c "
import paper_conf_icpp_lantra0m24_b200.build as b; b.build(force=True)" && echo "variants/libopp_$1.so"
