cd $GRAFT_REPO_ROOT
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python -m pytest tests -m gpu -x -q -k fused > gpurun_out/d3_pytest.log 2>&1
timeout 300 python scripts/ki2_producer.py > gpurun_out/d3_ki2.txt 2>&1
