#!/bin/bash
# Build experiment variants of libdgr in parallel (CPU): each variant reuses the
# product objects and recompiles only the listed sources with its -D flags.
#   tools/build_variants.sh NAME "DEFS" [NAME "DEFS" ...]
# -> paper_conf_sc_fernandonhzsgb22_b200/lib/libdgr_NAME.so (never the product)
set -e
cd "$(dirname "$0")/.."
PK=paper_conf_sc_fernandonhzsgb22_b200
python -c "from $PK import build as b; b.build()" > /dev/null
SRCS=${DGR_VARIANT_SRCS:-rhs_kernel.cu}
pids=()
while [ $# -ge 2 ]; do
  v=$1; d=$2; shift 2
  (
    od=$PK/lib/obj_$v; mkdir -p $od
    cp -p $PK/lib/obj/*.o $od/
    for s in $SRCS; do rm -f $od/${s//\//_}.o; done
    DGR_EXTRA_DEFS="$d" python -c "from $PK import build as b; b.build(variant='$v')" > /dev/null 2>$PK/lib/build_$v.log \
      && echo "built $v: $d" || { echo "FAILED $v"; cat $PK/lib/build_$v.log | tail -20; }
  ) &
  pids+=($!)
done
for p in "${pids[@]}"; do wait $p; done
