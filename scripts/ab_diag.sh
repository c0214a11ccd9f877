make host >/dev/null 2>&1
cp paper_conf_icpp_wrightdtcc23_b200/libnest.so /tmp/base.so
for v in base diagsm; do
  if [ $v = base ]; then cp /tmp/base.so paper_conf_icpp_wrightdtcc23_b200/libnest.so; else cp build_$v/libnest.so paper_conf_icpp_wrightdtcc23_b200/libnest.so; fi
  for spec in CFG2 G100; do echo "== $v $spec"; python scripts/ring_ab.py --spec $spec --configs quads --iters 5 2>&1 | grep -v "^{" | grep -v "S8"; done
done
cp /tmp/base.so paper_conf_icpp_wrightdtcc23_b200/libnest.so
