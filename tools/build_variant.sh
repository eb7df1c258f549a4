#!/bin/bash
# Build an A/B variant of libhdb: bash tools/build_variant.sh NAME "-DFOO=1 -DBAR=2"
# -> ab/libhdb_NAME.so (loaded by bench.py / tests through HDB_LIB=ab/libhdb_NAME.so)
cd "$(dirname "$0")/.."
NAME=$1; DEFS=$2
mkdir -p ab
make -s -C paper_conf_ipps_gowanlockrblp17_b200/csrc -j8 OUT=$PWD/ab/libhdb_$NAME.so BUILD=$PWD/ab/build_$NAME \
     NVFLAGS_EXTRA="$DEFS" CXXFLAGS_EXTRA="$DEFS" 2>&1 | grep -E "error|warning" ; ls -la ab/libhdb_$NAME.so
