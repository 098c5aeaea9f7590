python -c "import __graft_entry__ as g; g.build()" > gpurun_out/t_build.log 2>&1 || { tail -20 gpurun_out/t_build.log; exit 1; }
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3
timeout 2400 python -m pytest tests -m gpu -x -q ${1:+-k "$1"} > gpurun_out/t_pytest.log 2>&1; tail -5 gpurun_out/t_pytest.log
