set -u
mkdir -p gpurun_out
timeout 400 python tools/tts_run.py --workload random --n 32768 --fraction 0.9995 --also 0.99,0.995,0.999 --ref-seconds 60 --max-seconds 60 --repeats 3 > gpurun_out/tts_random32k.jsonl 2> gpurun_out/tts.err; echo "r32k rc=$?"
timeout 300 python tools/tts_run.py --workload random --n 1024 --fraction 1.0 --also 0.99,0.995,0.999 --ref-seconds 30 --max-seconds 30 --repeats 3 > gpurun_out/tts_random1k.jsonl 2>> gpurun_out/tts.err; echo "r1k rc=$?"
timeout 300 python tools/tts_run.py --workload maxcut --n 2000 --edges 19990 --fraction 1.0 --also 0.99,0.995,0.999 --ref-seconds 30 --max-seconds 30 --repeats 3 > gpurun_out/tts_maxcut2k.jsonl 2>> gpurun_out/tts.err; echo "mc rc=$?"
cat gpurun_out/tts_*.jsonl
