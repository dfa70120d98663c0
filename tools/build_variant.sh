#!/bin/bash
# Build libad from a source directory into ab/NAME.so (A/B variants; same flags as build.py):
#   bash tools/build_variant.sh NAME SRCDIR [extra nvcc flags...]
cd "$(dirname "$0")/.."
NAME=$1; SRC=$2; shift 2
FLAGS=$(python -c "from paper_conf_sc_solis_vasquezts25_b200 import build as B; print(' '.join(B.NVCC_FLAGS))")
mkdir -p ab
nvcc $FLAGS "$@" -I include -o ab/$NAME.so $SRC/ad_api.cu && echo ab/$NAME.so
