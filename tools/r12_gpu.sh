O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build.log 2>&1; echo build rc=$?
timeout 1200 python tools/reserve_ab.py --schedules overlap --reserves 0,32,128,512 > $O/reserve_ab2.jsonl 2> $O/reserve_ab2.err; echo ab rc=$?; cut -c1-330 $O/reserve_ab2.jsonl; tail -3 $O/reserve_ab2.err
mkdir -p $O/vs
timeout 300 python tools/vs_trace.py > $O/vs/trace.json 2> $O/vs/trace.err; echo trace rc=$?; tail -3 $O/vs/trace.err
