for L in pkg ab/st8.so; do
  LL=$L; [ "$L" = pkg ] && LL=$(pwd)/paper_conf_icde_giesekerhvo20_b200/libbfast.so
  echo "== $L"; BFAST_LIB=$LL timeout 300 python tools/periods_exp.py 2>&1 | grep "^{" | grep yearly7
done
