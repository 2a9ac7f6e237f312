bash tools/gpu/ab.sh "new sms4 sms10 sms16 sms33" 2
