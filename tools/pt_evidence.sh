o=gpurun_out/ptf
mkdir -p $o
timeout 900 python -m pytest tests/test_gpu_pt_forward.py -x -q > $o/tests.log 2>&1; echo rc=$? >> $o/tests.log
timeout 600 python tools/pt_transport_bench.py bert_base 128 10 > $o/pt_bert_base.jsonl 2> $o/pt_bert_base.err
timeout 600 python tools/pt_transport_bench.py bert_large 384 10 > $o/pt_bert_large.jsonl 2> $o/pt_bert_large.err
timeout 300 ncu --set full --clock-control none --import-source on -k regex:pt_forward -s 46 -c 1 -o $o/full_ptfwd -f python tools/kbench.py ptfwd 20 > $o/full_ptfwd.log 2>&1
ncu -i $o/full_ptfwd.ncu-rep --page raw --csv > $o/full_ptfwd.raw.csv 2>/dev/null
ncu -i $o/full_ptfwd.ncu-rep --page details --csv > $o/full_ptfwd.details.csv 2>/dev/null
timeout 120 python tools/kbench.py ptfwd 20 > $o/kbench_ptfwd.json 2>&1
