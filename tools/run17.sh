python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_new.py > gpurun_out/memcheck_new.log 2>&1; echo rc=$? >> gpurun_out/memcheck_new.log
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_case.py ip_f32_r4 > gpurun_out/racecheck_ip.log 2>&1; echo rc=$? >> gpurun_out/racecheck_ip.log
