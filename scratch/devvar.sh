#!/bin/bash
# usage: devvar.sh name "flags" [name "flags" ...]   (D=10 only builds)
cd /root/repo
while [ $# -gt 0 ]; do
  name=$1; flags=$2; shift 2
  EGG_OUT=scratch/variants/lib_$name.so EGG_BUILD_DIR=scratch/variants/build_$name EGG_NVCC_EXTRA="-DEGG_DEV_D=10 $flags" python paper_conf_edbt_jorgensena23_b200/build.py > scratch/variants/$name.log 2>&1 &
done
wait
