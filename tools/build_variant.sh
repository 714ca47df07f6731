# Build librtm from a git revision's csrc (or the working tree with "-") into the given .so path.
#   bash tools/build_variant.sh <rev|-> <out.so> [extra nvcc flags...]
REV=${1:?rev}; OUT=${2:?out}; shift 2
TMP=$(mktemp -d)
if [ "$REV" = "-" ]; then cp paper_conf_micro_mosallaeii024_b200/csrc/* $TMP/; cp include/rtm.h $TMP/;
else git show $REV:paper_conf_micro_mosallaeii024_b200/csrc/rtm_kernels.cu > $TMP/rtm_kernels.cu
     git show $REV:paper_conf_micro_mosallaeii024_b200/csrc/rtm_api.cpp > $TMP/rtm_api.cpp
     git show $REV:paper_conf_micro_mosallaeii024_b200/csrc/rtm_internal.h > $TMP/rtm_internal.h
     git show $REV:include/rtm.h > $TMP/rtm.h
     git show $REV:paper_conf_micro_mosallaeii024_b200/csrc/rtm_partition.cu > $TMP/rtm_partition.cu 2>/dev/null || rm -f $TMP/rtm_partition.cu; fi
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
  --expt-relaxed-constexpr -I $TMP "$@" -o $OUT $TMP/rtm_api.cpp $TMP/rtm_kernels.cu $( [ -f $TMP/rtm_partition.cu ] && echo $TMP/rtm_partition.cu ) && echo built $OUT
rm -rf $TMP
