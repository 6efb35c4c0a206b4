#!/bin/bash
# build encoder/decoder tuning variants (f32 ABS instantiations only) as libpfpl_<name>.so
# usage: tools/variants.sh name1 "-DFLAG=..." name2 "-DFLAG ..." ...
cd /root/repo
export PFPL_VARIANT_ONLY=${PFPL_VARIANT_ONLY:-enc_0_0,dec_0_0}
while [ $# -gt 1 ]; do
  n=$1; f=$2; shift 2
  python paper_conf_ipps_fallinadcb25_b200/_build.py libpfpl_$n.so $f > /tmp/var_$n.log 2>&1 && echo "built $n" || { echo "FAILED $n"; tail -5 /tmp/var_$n.log; }
done
