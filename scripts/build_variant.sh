#!/bin/bash
# build_variant.sh NAME "NVCC FLAGS": rebuild only the eval2 kernel translation
# units with extra flags and link abtest/lib_NAME.so against the in-tree objects
# of everything else (A/B and ablation timing via MAGIS_LIB).
set -e
name=$1; shift
flags="$*"
C=paper_conf_asplos_chend0zll024_b200/csrc
mkdir -p abtest/obj_$name
objs=""
for f in $C/*.o; do b=$(basename $f .o)
  case $b in magis_eval2_m*|magis_eval2_am) ;; *) objs="$objs $f";; esac
done
pids=""
for src in magis_eval2_m0t1 magis_eval2_m0t2 magis_eval2_m1 magis_eval2_m2 magis_eval2_m3 magis_eval2_am; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC -Xcompiler -fvisibility=hidden \
    --expt-relaxed-constexpr -I include -I $C -DMAGIS_BUILD $flags -c $C/$src.cu -o abtest/obj_$name/$src.o &
  pids="$pids $!"
done
for p in $pids; do wait $p; done
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o abtest/lib_$name.so $objs abtest/obj_$name/*.o -lcudart
echo abtest/lib_$name.so
