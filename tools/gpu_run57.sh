# initcheck re-run after the harness fix (sanitize_run.py copied the unwritten tail of the filter index buffer)
mkdir -p gpurun_out
timeout 900 compute-sanitizer --tool initcheck python tests/sanitize_run.py > gpurun_out/r57_initcheck.log 2>&1
echo done
