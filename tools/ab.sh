for v in libpfpl.so $VARS; do echo "== $v"; PFPL_LIB=$v timeout 300 python tools/bench_all.py $CASES 2>&1 | grep "^| [A-Z]" ; done
