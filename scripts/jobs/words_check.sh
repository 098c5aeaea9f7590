python -c "import __graft_entry__ as g; g.build()" > gpurun_out/w_build.log 2>&1 || { tail -20 gpurun_out/w_build.log; exit 1; }
timeout 600 python scripts/word_check.py c1 c2 c3 2>&1 | tail -20
