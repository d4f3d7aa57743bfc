cp paper_conf_sc_goldfarbjk13_b200/libtt.so /tmp/libtt_orig.so
for rep in 1 2 3; do for v in ${AB_LIBS:-base noself3}; do
  cp abtest/libtt_$v.so paper_conf_sc_goldfarbjk13_b200/libtt.so
  r=$(timeout 600 python bench.py --workload bhsteps --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(round(d['ms_per_step'],3))")
  echo "$v: $r"
done; done
cp /tmp/libtt_orig.so paper_conf_sc_goldfarbjk13_b200/libtt.so
