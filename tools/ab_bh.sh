rm -f gpurun_out/quick.jsonl
for i in 1 2; do
bash tools/quick_bench.sh "bh auto 10"
cp paper_conf_sc_goldfarbjk13_b200/libtt.so /tmp/libtt_base.so
cp libtt_gmem.so paper_conf_sc_goldfarbjk13_b200/libtt.so
bash tools/quick_bench.sh "bh auto 10"
cp /tmp/libtt_base.so paper_conf_sc_goldfarbjk13_b200/libtt.so
done
